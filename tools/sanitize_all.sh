#!/bin/bash
# compute-sanitizer over tools/sanitize_run.py, every tool; summaries to $1
out=${1:-gpurun_out/sanitizers.txt}
echo "# compute-sanitizer over tools/sanitize_run.py (every runtime mode x all 5 placements x fold, semantic programs 0-8, fork/join incl. one-warp teams, XS bucketed/plain/history/sorted/nuclide+hash grids/peer-combine epilogue, SU3 plain + GTR_F_TMA, RS wide+narrow poles), B200, $(date -u +%F)" > $out
for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
  echo "## $tool" >> $out
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py > /tmp/san_$tool.log 2>&1
  echo "rc=$?" >> $out
  grep -E "sanitize run ok|SUMMARY|Race reported|Warning|Error|hazard" /tmp/san_$tool.log | sed -E "s/\+0x[0-9a-f]+//" | sort | uniq -c | sort -rn | head -60 >> $out
done
