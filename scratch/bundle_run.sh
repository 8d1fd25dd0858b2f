# short-row bundles: GPU tests + A/B on C5
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/bundle_pytest.txt
run() {
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>gpurun_out/bundle_err_$p.txt | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>4}, d['clocks']['sm_mhz'])
" >> gpurun_out/bundle_ab.txt
  done
}
AGNN_SHORT_BUNDLES=0 run bundles=0
run bundles=1
AGNN_SHORT_BUNDLES=0 run bundles=0
run bundles=1
