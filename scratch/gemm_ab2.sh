LIB=paper_conf_sc_bestarglzcgssci23_b200/libagnn.so
timeout 900 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_training.py tests/test_gpu_multirank.py -q 2>&1 | tail -3 > gpurun_out/gemm2_pytest.txt
run() {
  cp scratch/libagnn_$1.so $LIB
  for c in C5 C4; do
    timeout 400 python bench.py --config $c --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$c', '$1', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if 'gemm' in k}, d['clocks']['sm_mhz'])
" >> gpurun_out/gemm_ab2.txt
  done
}
run head; run new; run head; run new
cp scratch/libagnn_new.so $LIB
