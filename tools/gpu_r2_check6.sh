# round-2 GPU check 6: mirrored execution + full GPU suite
set -x
timeout 900 python -m pytest tests/test_gpu_mirror.py -q -s -p no:cacheprovider -x > gpurun_out/r2_mirror.log 2>&1; echo "mirror rc=$?"
tail -30 gpurun_out/r2_mirror.log | grep -E "passed|failed|Error|error|assert" | head -20
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2_gputest8.log 2>&1; echo "pytest rc=$?"
grep -E "passed|failed" gpurun_out/r2_gputest8.log | tail -2; grep -E "^FAILED" gpurun_out/r2_gputest8.log | head
