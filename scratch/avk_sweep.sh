run() { python bench.py --config $1 --no-cpu-baseline --no-e2e --steps 5 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('%.3e'%d['value'], {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})"; }
for f in 0 1 2 3; do echo "fwd=$f"; AGNN_AVK_FWD=$f AGNN_AVK_BWD=0 run C3; done
for b in 1 2; do echo "bwd=$b"; AGNN_AVK_BWD=$b run C3; done
