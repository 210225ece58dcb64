#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_peer_exchange_gpu.py tests/test_dist_nccl_gpu.py -x -q 2>&1 | tail -25 > gpurun_out/r02c_tests.txt
python - > gpurun_out/r02c_mc.txt 2>&1 <<'PY'
from cuda.bindings import driver as d
d.cuInit(0)
err, dev = d.cuDeviceGet(0)
for name in ("CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED", "CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED",
             "CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR_SUPPORTED"):
    a = getattr(d.CUdevice_attribute, name, None)
    print(name, d.cuDeviceGetAttribute(a, dev) if a is not None else "n/a")
PY
cat gpurun_out/r02c_tests.txt gpurun_out/r02c_mc.txt
