mkdir -p gpurun_out
for cfg in "" "-DPEPP_Y_EVICT_FIRST=1"; do
  PEPP_NVCC_EXTRA="$cfg" python build.py --force > /dev/null 2>&1 || echo build_failed
  echo "== $cfg"; timeout 900 python tools/r2/wl_time.py uniform1m zipf4m 2>&1 | grep '^{'; timeout 900 python tools/r2/panel_mid.py 10000000 12000000 16000000 2>&1 | grep '^{' | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print(d['rows'], d['us'].get('sell[1]'), d['us'].get('csr_vector[8]'), d['us'].get('panel[22]'))"
done
