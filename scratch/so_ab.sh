# A/B of two builds of libagnn.so (scratch/libagnn_head.so vs scratch/libagnn_new.so) on C5
LIB=paper_conf_sc_bestarglzcgssci23_b200/libagnn.so
run() {
  cp scratch/libagnn_$1.so $LIB
  for p in fp32 bf16; do
    timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', '$1', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>4}, d['clocks']['sm_mhz'])
" >> gpurun_out/so_ab.txt
  done
}
run head; run new; run head; run new
cp scratch/libagnn_new.so $LIB
