set -u
O=gpurun_out/r2p; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_records -s 4 -c 1 -o $O/full_s1 python bench.py --config s1 --steps 1 --warmup 4 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo "full s1 rc=$?"
TAG=r2p/storm CFGS="s1 s2 c2" bash tools/storm_ncu.sh
TAG=r2p/storm_noagg CFGS="s1 s2" BENCH_ARGS="--no-warp-agg" bash tools/storm_ncu.sh
