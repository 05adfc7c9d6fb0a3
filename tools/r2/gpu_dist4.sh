# reproduce: 4-rank distribution test (fake NCCL, one GPU), default build vs single-line pattern tiles
mkdir -p gpurun_out
for cfg in "" "-DPEPP_MTILE_K=1" "-DPEPP_PTILE=0"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || { echo build_failed; continue; }
  echo "== $cfg"
  timeout 400 python -m pytest tests/test_gpu_partitioned.py -q -p no:cacheprovider -x -k "distribution_choice_agreed_and_bitwise and lap-4" --timeout 300 > gpurun_out/dist4.log 2>&1; echo rc=$?; tail -2 gpurun_out/dist4.log
  nvidia-smi --query-gpu=utilization.gpu --format=csv,noheader
done
