# BF16 storage mode: GPU tests, bench (default + MINB variants), ncu launch list
set -x
timeout 600 python -m pytest tests/test_gpu_bf16.py -q 2>&1 | tail -25 > gpurun_out/pytest_bf16.txt
timeout 300 python bench.py --prec bf16 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_bf16.json 2> gpurun_out/bench_c5_bf16.err
AGNN_BWD_MINB=3 timeout 300 python bench.py --prec bf16 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_bf16_b3.json 2>&1
AGNN_FWD_MINB=4 timeout 300 python bench.py --prec bf16 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_bf16_f4.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
   --log-file gpurun_out/r01_launches_c5_bf16.csv \
   python bench.py --prec bf16 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench_c5_bf16.log 2>&1
