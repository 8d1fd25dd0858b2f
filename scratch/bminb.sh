run() {
    timeout 300 python bench.py --prec fp32 --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('fp32', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if 'short' in k}, d['clocks']['sm_mhz'])
" >> gpurun_out/bminb.txt
}
run base; AGNN_BUNDLE_MINB=3 run minb3; run base; AGNN_BUNDLE_MINB=3 run minb3
