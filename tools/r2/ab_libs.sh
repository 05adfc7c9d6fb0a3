# A/B of library builds (tools/r2/libs/*.so) on one command: each build is copied in place, the command runs twice
cmd="$1"
for rep in 1 2; do
for lib in tools/r2/libs/*.so; do
  cp $lib paper_conf_sc_dastgeerlk12_b200/libpepp_spmv.so
  echo "== $lib (rep $rep)"; eval "$cmd"
done; done
