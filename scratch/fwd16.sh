timeout 900 python -m pytest tests/test_gpu_bf16.py tests/test_gpu_factored.py -q 2>&1 | tail -3 > gpurun_out/fwd16_pytest.txt
run() {
    timeout 300 python bench.py --prec bf16 --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('bf16', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if 'fwd' in k}, d['clocks']['sm_mhz'])
" >> gpurun_out/fwd16.txt
}
for v in 1 0 2 1 0; do AGNN_FWD16_VARIANT=$v run v=$v; done
