#!/bin/bash
# full GPU test suite + smoke; logs under gpurun_out/$1
O=gpurun_out/${1:-tests}; mkdir -p $O
timeout 300 python __graft_entry__.py smoke > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 ${PYTEST_ARGS} > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
tail -3 $O/smoke.log; grep -E "passed|failed|error" $O/pytest_gpu.log | tail -5
