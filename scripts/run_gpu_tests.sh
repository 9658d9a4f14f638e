#!/bin/bash
# helper for gpurun: smoke, GPU tests, short bench
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5
timeout ${TEST_TIMEOUT:-1200} python -m pytest tests -m gpu -q --timeout 900 ${PYTEST_ARGS} 2>&1 | tail -40 > gpurun_out/pytest_gpu.txt
tail -40 gpurun_out/pytest_gpu.txt
