# session 3: sanitizer passes over the new kernels (block spans, replicated ring, host pipeline)
mkdir -p gpurun_out
( echo "== memcheck: block spans, random types, every kernel family (small), record spans"
  timeout 1200 compute-sanitizer --tool memcheck --leak-check no python -m pytest tests/test_gpu_parity.py -q -k "block_span or random or (every_kernel and not C2s) or record_span" 2>&1 | tail -3
  echo "== racecheck: block spans (pack+unpack, smem maps and TMA windows)"
  timeout 900 compute-sanitizer --tool racecheck python -m pytest tests/test_gpu_parity.py -q -k "block_span and (shuffled4 or gran8 or jumps4)" 2>&1 | tail -3
  echo "== synccheck: block spans"
  timeout 900 compute-sanitizer --tool synccheck python -m pytest tests/test_gpu_parity.py -q -k "block_span and (shuffled4 or descending)" 2>&1 | tail -3
  echo "== memcheck: ring with replicas and block spans"
  timeout 900 compute-sanitizer --tool memcheck --leak-check no python -m pytest tests/test_gpu_xfer.py -q -k "replicas or block_spans" 2>&1 | tail -3
) > gpurun_out/sanitizer_s3.txt 2>&1
cat gpurun_out/sanitizer_s3.txt
