# DSMEM gather probe (tools/experiments/dsmem_probe.cu)
mkdir -p gpurun_out
cd tools/experiments && timeout 300 ./dsmem_probe > ../../gpurun_out/dsmem_probe.log 2>&1; echo probe_rc=$?; cat ../../gpurun_out/dsmem_probe.log
