cd "${GRAFT_REPO_ROOT:-/root/repo}"
O=gpurun_out/r02i; mkdir -p $O
(cd build/oldtree && timeout 300 python tools/time_kmeans.py > ../../$O/old_time.log 2>&1)
timeout 300 python tools/time_kmeans.py > $O/new_time.log 2>&1
(cd build/oldtree && timeout 900 ncu --set full --import-source on --clock-control none -k regex:kmeans_tma -s 2 -c 1 -o ../../$O/old_km python tools/profile_items.py kmeans > ../../$O/old_ncu.log 2>&1)
timeout 900 ncu --set full --import-source on --clock-control none -k regex:kmeans_tma -s 2 -c 1 -o $O/new_km python tools/profile_items.py kmeans > $O/new_ncu.log 2>&1
ls $O
