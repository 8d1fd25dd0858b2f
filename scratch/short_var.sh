# short-row kernel variants (factored path), C5 fp32 + bf16
run() {
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if 'short' in k}, d['clocks']['sm_mhz'])
" >> gpurun_out/short_var.txt
  done
}
run base
for v in 1 2; do AGNN_FWD_SHORT_VARIANT=$v AGNN_BWD_SHORT_VARIANT=$v run v=$v; done
AGNN_BWD_SHORT_VARIANT=3 run bwd=3
run base
