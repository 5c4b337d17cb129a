#!/bin/bash
# full GPU suite with the full-size cfg4 growth test
OUT=gpurun_out/r3u; mkdir -p $OUT
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/gpu_tests.log 2>&1; tail -3 $OUT/gpu_tests.log
grep -n "cfg4_full" $OUT/gpu_tests.log | head -3
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k cfg4_full --durations=3 > $OUT/cfg4_test.log 2>&1; tail -6 $OUT/cfg4_test.log
