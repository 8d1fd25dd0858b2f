# quick kernel-time comparison: bench.py bf16 and fp32 C5, 5 steps
for p in ${PRECS:-bf16 fp32}; do
  timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p ${TAG:-}', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})
"
done
