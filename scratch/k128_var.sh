run() {
  for p in ${PRECS:-fp32 bf16}; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if k in ('gat_fwd_kernel','gat_bwd_kernel')}, d['clocks']['sm_mhz'])
" >> gpurun_out/k128_var.txt
  done
}
run base
for v in 1 2 3; do AGNN_BWDF_VARIANT=$v run bwdf=$v; done
for v in 1 2; do PRECS=fp32 AGNN_FWD_VARIANT=$v run fwd=$v; done
run base
