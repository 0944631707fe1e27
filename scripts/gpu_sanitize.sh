#!/bin/bash
# compute-sanitizer over scripts/sanitize_case.py (every kernel variant, small inputs)
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  extra=""
  # NCCL's ncclMemAlloc probes cuMemCreate handle types and falls back when one is refused; the
  # refused probe is a host API error inside libnccl, not a device fault, so memcheck reports
  # device-side errors only (--report-api-errors no); the API error is logged by the first pass
  if [ $tool = memcheck ]; then
    timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python scripts/sanitize_case.py > gpurun_out/sanitize_memcheck_api.log 2>&1
    echo "memcheck (API errors reported) rc=$?"; grep -E "Program hit|SUMMARY" gpurun_out/sanitize_memcheck_api.log
    extra="--report-api-errors no"
  fi
  timeout 900 compute-sanitizer --tool $tool $extra --print-limit 20 --error-exitcode 9 python scripts/sanitize_case.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -2 gpurun_out/sanitize_$tool.log
done
