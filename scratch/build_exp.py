"""Build experiment variants of libagnn.so: python scratch/build_exp.py tag DEF1 DEF2 ..."""
import sys
sys.path.insert(0, "/root/repo")
from paper_conf_sc_bestarglzcgssci23_b200 import _build
tag, defs = sys.argv[1], sys.argv[2:]
print(_build.build_agnn(force=True, out=f"/root/repo/scratch/libagnn_{tag}.so", defines=defs))
