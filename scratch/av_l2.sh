timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_training.py tests/test_gpu_multirank.py -q 2>&1 | tail -3 > gpurun_out/av_pytest.txt
run() {
  for c in C4 C3; do
    timeout 400 python bench.py --config $c --steps 5 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$c', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1}, d['clocks']['sm_mhz'])
" >> gpurun_out/av_l2.txt
  done
}
AGNN_L2_HOT_MB=0 run hot=0
run hot=96
AGNN_L2_HOT_MB=0 run hot=0
run hot=96
