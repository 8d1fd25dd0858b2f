timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_factored.py -q -x 2>&1 | tail -3 > gpurun_out/xw_pytest.txt
run() {
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if k in ('gat_fwd_kernel','gat_bwd_kernel')}, d['clocks']['sm_mhz'])
" >> gpurun_out/xw_ab.txt
  done
}
AGNN_XW_PREFETCH=0 run xw=0; run xw=1; AGNN_XW_PREFETCH=0 run xw=0; run xw=1
