# A/B timing of library variants via env: AB_SPECS="C2 0.5|C2 4" bash tools/ab.sh TAG "ENV1" "ENV2" ...
TAG=$1; shift
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || exit 1
: > gpurun_out/ab_$TAG.jsonl
IFS='|' read -ra SPECS <<< "${AB_SPECS:-C2 0.5|C2 4}"
for envs in "$@"; do
  for spec in "${SPECS[@]}"; do
    set -- $spec
    out=$(env $envs timeout 600 python tools/time_job.py $1 $2 ${3:-1} 2>&1 | tail -1)
    echo "{\"env\": \"$envs\", \"spec\": \"$spec\", \"r\": $out}" >> gpurun_out/ab_$TAG.jsonl
  done
done
