# quality tests + sanitizers on the r02 kernels (summaries -> gpurun_out/san/summary.txt)
mkdir -p gpurun_out/san
timeout 900 python -m pytest tests/test_gpu_quality.py -m gpu -q -p no:cacheprovider 2>&1 | tail -5 > gpurun_out/pytest_quality.txt
for c in lean_c1 lean_c4s lean_c4s_fp32 lean_c2 shards general_c4s step_c4s step_16b infer sparse; do
  for tool in memcheck racecheck synccheck; do
    extra=""; [ $tool = racecheck ] && extra="--racecheck-report hazard"
    timeout 600 compute-sanitizer --tool $tool $extra --print-limit 200 python tools/sanitize_cases.py $c > gpurun_out/san/${c}_${tool}.txt 2>&1
    echo "$c $tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san/${c}_${tool}.txt | tail -1) $(grep -c 'case .* ok' gpurun_out/san/${c}_${tool}.txt) parity-ok" >> gpurun_out/san/summary.txt
  done
done
timeout 900 compute-sanitizer --tool memcheck --target-processes all python -m pytest tests/test_gpu_sharding.py -q -p no:cacheprovider -k two_processes > gpurun_out/san/ipc_memcheck.txt 2>&1
echo "ipc_two_processes memcheck rc=$? $(grep -E 'ERROR SUMMARY' gpurun_out/san/ipc_memcheck.txt | tail -2 | tr '\n' ' ') $(grep -E 'passed|failed' gpurun_out/san/ipc_memcheck.txt | tail -1)" >> gpurun_out/san/summary.txt
cat gpurun_out/pytest_quality.txt; cat gpurun_out/san/summary.txt
