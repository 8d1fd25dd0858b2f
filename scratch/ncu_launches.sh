# launch list (+ DRAM bytes) of one bench step per config, ncu serialised, cold cache
for c in C5 C3 C4; do
  ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
      --log-file gpurun_out/r01_launches_$(echo $c | tr A-Z a-z).csv \
      python bench.py --config $c --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench_$c.log 2>&1
done
ls -la gpurun_out/
