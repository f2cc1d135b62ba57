# A/B timing of the raw-text job: bash tools/ab_text.sh TAG "ENV1" "ENV2" ...  (ratios: AB_RATIOS, default "4 0.5")
TAG=$1; shift
: > gpurun_out/abt_$TAG.jsonl
for envs in "$@"; do
  env $envs timeout 600 python tools/time_text.py ${AB_RATIOS:-4 0.5} 2>&1 | grep '^{' | sed "s/^/{\"env\": \"$envs\", \"r\": /; s/$/}/" >> gpurun_out/abt_$TAG.jsonl
done
