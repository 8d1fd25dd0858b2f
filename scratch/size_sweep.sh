# C5 recipe (GAT, Kronecker ef 32, k = 128, 4 heads) at n = 2^21 .. 2^24 on one GPU:
# the per-GPU points of the weak-scaling series n_P = 2^21 P
for sc in 21 22 23 24; do
  timeout 400 python bench.py --scale $sc --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
r=d['roofline']
print('n=2^$sc', 'edges', d['config']['edges'], 'edges/s %.3e' % d['value'], 'ms/step %.2f' % d['ms_per_step'], 'dominant', r['pass'], 'model frac %.2f' % r['model_frac'], 'clock', d['clocks']['sm_mhz'])
" >> gpurun_out/r02_size_sweep.txt
done
