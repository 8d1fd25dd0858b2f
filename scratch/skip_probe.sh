# time the sparse kernels with short rows removed from the work list (debug knob)
for d in 0 4 16 64 2049; do
  for p in bf16 fp32; do
  AGNN_DEBUG_SKIP_BELOW=$d timeout 300 python bench.py --prec $p --steps 3 --warmup 2 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
k=d['kernels']
print('skip<$d $p', 'fwd', round(k['gat_fwd_kernel']['ms_per_step'],2), 'bwd', round(k['gat_bwd_kernel']['ms_per_step'],2))
" >> gpurun_out/skip_probe.txt
  done
done
cat gpurun_out/skip_probe.txt
