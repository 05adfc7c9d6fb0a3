# value compression: parity + bench on / off + ncu traffic of the compressed SELL kernel
mkdir -p gpurun_out
python build.py > /dev/null
python -m pytest tests/test_gpu_parity.py tests/test_gpu_fp32.py tests/test_gpu_fullsize.py -x -q 2>&1 | tail -3
python bench.py --no-cpu --no-sweep 2>/dev/null | tail -1 > gpurun_out/vc_on.json
python bench.py --no-cpu --no-sweep --no-value-compression 2>/dev/null | tail -1 > gpurun_out/vc_off.json
python -c "
import json
for f in ['on','off']:
    d=json.load(open('gpurun_out/vc_%s.json'%f)); print(f, d['value'], d['roofline']['avg_launch_us'], d['roofline']['kernel'], d['plan']['sell_constval_frac'], d['e2e']['value'])"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"sell_kernel" -c 1 -o gpurun_out/prof_sell_lap_vc python tools/prof_run.py --workload lap8192 --variants sell --reps 1 > gpurun_out/ncu_vc.log 2>&1; echo ncu=$?
