#!/bin/bash
set -u
O=gpurun_out
mkdir -p $O
timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python -m pytest tests/test_gpu_fuzz.py -q -x -k "test_fuzz_case and (8 or 9)" > $O/san_fuzz8_r02l.log 2>&1
timeout 600 python -m pytest tests/test_gpu_fuzz.py -q -x > $O/fuzz_r02l.log 2>&1
echo done
