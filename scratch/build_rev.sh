#!/bin/bash
# build libagnn.so of git revision $1 into scratch/libagnn_$2.so (A/B timing with AGNN_LIB)
set -e
rev=$1; tag=$2
d=$(mktemp -d)
git -C /root/repo archive $rev | tar -x -C $d
cd $d && python -c "
import sys; sys.path.insert(0, '.')
from paper_conf_sc_bestarglzcgssci23_b200 import _build; _build.build_agnn(force=True)" > /dev/null 2>&1
cp $d/paper_conf_sc_bestarglzcgssci23_b200/libagnn.so /root/repo/scratch/libagnn_$tag.so
rm -rf $d
echo built scratch/libagnn_$tag.so
