# L2 residency hints: budget sweep on C5 (fp32, bf16), hot=0 bracketing for drift
run() {
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>5}, d['clocks']['sm_mhz'])
" >> gpurun_out/l2_sweep2.txt
  done
}
AGNN_L2_HOT_MB=0 run hot=0
for b in 64 128 192 256 400; do AGNN_L2_HOT_MB=$b run hot=$b; done
AGNN_L2_HOT_MB=0 run hot=0
