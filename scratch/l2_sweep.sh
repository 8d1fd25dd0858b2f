# L2 residency hints sweep on C5 (fp32 and bf16): budget MB x cold policy x set-aside
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bf16.py -x -q 2>&1 | tail -3 > gpurun_out/l2_pytest.txt
run() {
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})
" >> gpurun_out/l2_sweep.txt
  done
}
AGNN_L2_HOT_MB=0 run hot=0
AGNN_L2_HOT_MB=64 run hot=64 cold=first
AGNN_L2_HOT_MB=64 AGNN_L2_COLD=0 run hot=64 cold=normal
AGNN_L2_HOT_MB=32 run hot=32
AGNN_L2_HOT_MB=100 run hot=100
AGNN_L2_HOT_MB=64 AGNN_L2_SETASIDE_MB=80 run hot=64 setaside=80
AGNN_L2_HOT_MB=100000 AGNN_L2_COLD=0 run hot=all-last
