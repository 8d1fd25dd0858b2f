timeout 1200 python -m pytest tests/test_gpu_factored.py tests/test_gpu_parity.py tests/test_gpu_training.py tests/test_gpu_multirank.py -q 2>&1 | tail -6 > gpurun_out/genfact_pytest.txt
run() {
    timeout 300 python bench.py --config C2 --steps 20 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('C2', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k:round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.02})
" >> gpurun_out/genfact_ab.txt
}
AGNN_GAT_FACTORED=0 run fac=0; run fac=1; AGNN_GAT_FACTORED=0 run fac=0; run fac=1
