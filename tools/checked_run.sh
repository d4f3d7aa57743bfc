#!/bin/bash
# Checked build (build.py --checked: device-side bounds checks, tt_check.cuh)
# over the whole GPU test suite and the sanitizer workload (every kernel,
# variant and mode) -- the stand-in for compute-sanitizer, which this pool
# has closed.  Logs in gpurun_out/checked/.
mkdir -p gpurun_out/checked
python -c "import sys; sys.path.insert(0, '.'); import paper_conf_sc_goldfarbjk13_b200.build as B; print(B.build(checked=True))" > gpurun_out/checked/build.txt 2>&1
TT_LIB=checked timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/checked/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> gpurun_out/checked/pytest_gpu.txt
TT_LIB=checked timeout 600 python tools/sanitize.py > gpurun_out/checked/sanitize_workload.txt 2>&1
echo "sanitize workload rc=$?" >> gpurun_out/checked/sanitize_workload.txt
TT_LIB=checked python -c "import paper_conf_sc_goldfarbjk13_b200._lib as L; print('loaded', L.LIB_PATH)" >> gpurun_out/checked/build.txt 2>&1
tail -2 gpurun_out/checked/pytest_gpu.txt; tail -3 gpurun_out/checked/sanitize_workload.txt
