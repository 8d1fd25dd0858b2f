# L2 hint budget sweep (fine classes) on C5, factored path
timeout 600 python -m pytest tests/test_gpu_factored.py -q -x 2>&1 | tail -3 > gpurun_out/l2s3_pytest.txt
run() {
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>5}, d['clocks']['sm_mhz'])
" >> gpurun_out/l2_sweep3.txt
  done
}
for b in 0 48 64 80 96 112 128 0; do AGNN_L2_HOT_MB=$b run hot=$b; done
