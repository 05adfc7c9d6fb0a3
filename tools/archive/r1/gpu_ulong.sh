# fp64 stencil list, offset sets of 9-16 slots (banded b = 4): U_LONG = 6 / 8 / 10 / 12, two repeats (alternating builds)
mkdir -p gpurun_out
for rep in 1 2; do
for u in 6 8 10 12; do
  PEPP_NVCC_EXTRA="-DPEPP_SLIST_U_F64_LONG=$u" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python tools/banded_ab.py --rows 1e7,1e8 2>&1 | grep banded | sed "s/^/U_long=$u /" | cut -c1-90
done
done
python build.py --force > /dev/null 2>&1
