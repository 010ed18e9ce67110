#!/bin/bash
# A/B of prebuilt libdgr variants + one ncu capture of the KBF launch of the first (usage: scratch/ab_run.sh TAG lib...)
TAG=$1; shift
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail $O/build.log; exit 1; }
scratch/ab.sh "$@" 2>&1 | tee $O/ab.txt
DGR_LIB=$1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:tile_bulk -s 3 -c 1 -o $O/kbf python tools/prof_run.py ispd19 3 > $O/ncu.log 2>&1
python tools/ncu_summary.py $O/kbf.ncu-rep 2>&1 | tee $O/ncu_summary.txt
