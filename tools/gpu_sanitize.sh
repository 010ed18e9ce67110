#!/bin/bash
# compute-sanitizer on the final kernels: memcheck / racecheck / synccheck / initcheck over tools/san_run.py
# usage: tools/gpu_sanitize.sh TAG
O=gpurun_out/${1:-san}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
run() {   # tool config [env...]
  local tool=$1 cfg=$2 tag=$3; shift 3
  env "$@" timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/san_run.py $cfg > $O/san_${tool}_${tag}.log 2>&1
  echo "== san_${tool}_${tag} (rc=$?)"; grep -E "san_run ok|ERROR SUMMARY|RACECHECK SUMMARY" $O/san_${tool}_${tag}.log | tail -2
}
for tool in memcheck racecheck synccheck initcheck; do
  run $tool tiny tiny
  run $tool c1e4 c1e4
  run $tool tiny_m tiny_m
done
run memcheck c1e4 c1e4_tiles32 DGR_TILE_BUNDLES=32
run racecheck c1e4 c1e4_tiles32 DGR_TILE_BUNDLES=32
run memcheck c1e4 c1e4_slow DGR_ALL_SLOW=1
run racecheck c1e4 c1e4_slow DGR_ALL_SLOW=1
