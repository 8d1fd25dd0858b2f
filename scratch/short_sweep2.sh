# short-row threshold sweep with the factored kernels (C5, fp32 + bf16)
run() {
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>5}, d['clocks']['sm_mhz'])
" >> gpurun_out/short_sweep2.txt
  done
}
for t in 32 0 4 8 16 32; do AGNN_SHORT_EDGES=$t run short=$t; done
