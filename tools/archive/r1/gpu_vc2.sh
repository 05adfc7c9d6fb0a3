mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "compression or hybrid or every_variant" > gpurun_out/pytest_vc2.log 2>&1; echo pytest_rc=$?; tail -3 gpurun_out/pytest_vc2.log
timeout 600 python bench.py --no-cpu --no-sweep --no-library --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.load(sys.stdin); print('headline', d['roofline']['avg_launch_us'], 'vc', d['value_compressed']['avg_launch_us'], d['value_compressed'].get('traffic_frac'), d['clocks']['sm_mhz'])"
