#!/bin/bash
# compute-sanitizer pass over the CUDA path (memcheck / racecheck / synccheck / initcheck).
# Run on a GPU box from the repo root:  bash tools/sanitize.sh [outdir]
# The torch caching allocator is disabled so every library allocation is its own cudaMalloc
# and memcheck sees the true bounds of each buffer.
out=${1:-gpurun_out/sanitize}
mkdir -p "$out"
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
CS="compute-sanitizer --print-limit 20 --error-exitcode 99"
SMOKE='import __graft_entry__ as g; g.smoke()'
for tool in memcheck racecheck synccheck initcheck; do
  timeout 600 $CS --tool $tool python -c "$SMOKE" > "$out/smoke_$tool.log" 2>&1
  echo "smoke $tool rc=$?" >> "$out/summary.txt"
done
# small-size parity tests (full-size and config-3 cases excluded: the sanitizer slows kernels ~100x)
for f in test_gpu_convert test_gpu_spmv test_gpu_spgemm test_gpu_vcycle test_gpu_pcg test_gpu_interp test_gpu_pmis test_gpu_dist; do
  timeout 900 $CS --tool memcheck python -m pytest tests/$f.py -m gpu -q -x -p no:cacheprovider \
      -k "not full and not cfg" > "$out/${f}_memcheck.log" 2>&1
  echo "$f memcheck rc=$? $(grep -h -E '^[0-9]+ (passed|failed)|passed|ERROR SUMMARY' "$out/${f}_memcheck.log" | tail -2 | tr '\n' ' ')" >> "$out/summary.txt"
done
# shared-memory races in the kernels with intra-CTA communication (A*P numeric's cp.async B
# staging and shared C rows, the symbolic kernels, the tail kernel): racecheck on small cases
for f in test_gpu_vcycle test_gpu_spgemm; do
  timeout 1200 $CS --tool racecheck python -m pytest tests/$f.py -m gpu -q -x -p no:cacheprovider \
      -k "not full and not cfg and not long" > "$out/${f}_racecheck.log" 2>&1
  echo "$f racecheck rc=$? $(grep -h -E 'passed|ERROR SUMMARY' "$out/${f}_racecheck.log" | tail -2 | tr '\n' ' ')" >> "$out/summary.txt"
done
grep -h "ERROR SUMMARY" "$out"/*.log | sort | uniq -c >> "$out/summary.txt"
