# banded b = 4 SELL time: paired-chunk build on / off
mkdir -p gpurun_out
for p in 0 1; do
  PEPP_NVCC_EXTRA="-DPEPP_SELL_PAIR_F64=$p" python build.py --force > /dev/null 2>&1 || echo build failed
  timeout 600 python tools/banded_ab.py --rows 1e7,1e8 2>&1 | sed "s/^/pair=$p /" | grep banded
done
python build.py --force > /dev/null 2>&1
