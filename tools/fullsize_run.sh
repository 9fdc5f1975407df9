#!/bin/bash
# One-off full-size parity sets of SURVEY §8(d) against the oracle (about 35 minutes of
# host-core oracle time): run under gpurun, the log lands in gpurun_out/fullsize.txt.
O=${1:-gpurun_out}; mkdir -p $O
{ echo "# Full-size parity sets of SURVEY §8(d) vs the oracle (SMILER_FULLSIZE=1 pytest tests/test_gpu_fullsize.py -m gpu -v -s),"
  echo "# one B200 + the box's $(nproc) host cores ($(grep -m1 'model name' /proc/cpuinfo)), code at commit $(cat .git_head 2>/dev/null || echo unknown)"
  SMILER_FULLSIZE=1 timeout 3300 python -m pytest tests/test_gpu_fullsize.py -m gpu -v -s -p no:cacheprovider 2>&1; } > $O/fullsize.txt
tail -3 $O/fullsize.txt
