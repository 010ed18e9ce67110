#!/bin/bash
# same-box A/B of libdgr variants (tools/ab_time.py); usage: tools/gpu_ab.sh TAG CONFIG lib1.so [lib2.so ...]
TAG=$1; CFG=$2; shift 2
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for round in 1 2; do
  for lib in "$@"; do
    if [ "$lib" = default ]; then python tools/ab_time.py $CFG 200 3; 
    elif [ "$lib" = kgcta ]; then DGR_KG_CTA=1 python tools/ab_time.py $CFG 200 3;
    else DGR_LIB=$PWD/$lib python tools/ab_time.py $CFG 200 3; fi
  done
done 2>&1 | grep -v Warning | tee $O/ab.jsonl
