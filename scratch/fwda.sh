AGNN_FWD_VARIANT=4 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gat or inference" 2>&1 | tail -3 > gpurun_out/fwda_pytest.txt
run() {
    timeout 300 python bench.py --prec fp32 --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>gpurun_out/fwda_err.txt | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('fp32', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if k in ('gat_fwd_kernel','gat_bwd_kernel')}, d['clocks']['sm_mhz'])
" >> gpurun_out/fwda.txt
}
run base; AGNN_FWD_VARIANT=4 run v4; AGNN_FWD_VARIANT=5 run v5; run base; AGNN_FWD_VARIANT=4 run v4
