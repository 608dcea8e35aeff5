set -u
O=gpurun_out/r2h; mkdir -p $O
python __graft_entry__.py build > $O/build.log 2>&1 || { tail -30 $O/build.log; exit 1; }
timeout 600 python tools/warp_times.py c3 c2 > $O/wt_cur.txt 2>&1; grep -E "^c[0-9]" $O/wt_cur.txt
WT_SRC=$PWD/build/r1src WT_TAG=_r1 timeout 600 python tools/warp_times.py c3 c2 > $O/wt_r1.txt 2>&1; grep -E "^c[0-9]" $O/wt_r1.txt
