# ncu --set full of the factored GAT kernels at C5 (fp32 and bf16) + quick A/B
timeout 900 python -m pytest tests/test_gpu_factored.py tests/test_gpu_parity.py -q -x 2>&1 | tail -5 > gpurun_out/fact_pytest3.txt
for p in fp32 bf16; do
  timeout 300 python bench.py --prec $p --steps 5 --no-cpu-baseline --no-e2e --no-bf16-line 2>/dev/null | python -c "
import json,sys
d=json.loads([l for l in sys.stdin if l.startswith('{')][-1])
print('$p', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1}, d['clocks']['sm_mhz'])
" >> gpurun_out/fact_ab3.txt
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"gat_fwd_k128|gat_bwd_k128f|gat_fwd_short|gat_bwd_short" -c 4 \
     -o gpurun_out/fact_$p python bench.py --prec $p --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-bf16-line > gpurun_out/ncu_fact_$p.log 2>&1
done
