mkdir -p gpurun_out
echo "== default"; timeout 900 python tools/r2/wl_time.py zipf4m skew uniform1m 2>&1 | grep '^{'
PEPP_NVCC_EXTRA="-DPEPP_SELL_PAIR_SORTED=1" python build.py --force > /dev/null 2>&1 || echo build_failed
echo "== pair sorted"; timeout 900 python tools/r2/wl_time.py zipf4m skew uniform1m 2>&1 | grep '^{'
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -p no:cacheprovider -k "zipf or skew or config3" > gpurun_out/pairsorted_pytest.log 2>&1; echo pytest_rc=$?; tail -1 gpurun_out/pairsorted_pytest.log
