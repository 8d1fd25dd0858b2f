# final round validation: GPU tests, smoke, C5 ncu launch lists, default bench, reference arm
set -x
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -15 > gpurun_out/final_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.txt 2>&1
CONFIGS=C5 PRECS="fp32 bf16" bash scratch/ncu_launches.sh
timeout 600 python bench.py > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_ref.json 2> gpurun_out/final_ref.err
