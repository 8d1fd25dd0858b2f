# GEMM restructure: GEMM parity tests + per-kernel times at C5 / C4
timeout 900 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_training.py tests/test_gpu_multirank.py -q 2>&1 | tail -3 > gpurun_out/gemm_pytest.txt
for c in C5 C4; do
  timeout 400 python bench.py --config $c --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>gpurun_out/gemm_err.txt | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$c', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if 'gemm' in k}, d['clocks']['sm_mhz'])
" >> gpurun_out/gemm_ab.txt
done
