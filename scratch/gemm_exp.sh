export PYTHONPATH=$PWD
for e in 0 1 2 4 3 5 6 7; do echo "exp=$e"; AGNN_GEMM_EXP=$e python -c "
import sys; sys.argv=['x']
exec(open('scratch/gemm_probe.py').read().split('if __name__')[0])
timing(1<<24,128,144); timing(1<<24,128,128)"; done
