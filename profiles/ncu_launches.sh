# launch list (+ DRAM bytes) of one bench step per config, ncu serialised, cold cache
for c in ${CONFIGS:-C5 C3 C4}; do
  for p in ${PRECS:-fp32}; do
  tag=$(echo $c | tr A-Z a-z)$( [ $p = fp32 ] || echo _$p )
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
      --log-file gpurun_out/${ROUND:-r02}_launches_$tag.csv \
      python bench.py --config $c --prec $p --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-bf16-line > gpurun_out/ncu_bench_$tag.log 2>&1
  done
done
ls -la gpurun_out/
