#!/bin/bash
# the GPU suite twice back to back (flakiness check) + smoke
mkdir -p gpurun_out
for i in 1 2; do timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/flaky_$i.log 2>&1; echo "rc=$?" >> gpurun_out/flaky_$i.log; done
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke2.log 2>&1; echo "rc=$?" >> gpurun_out/smoke2.log
