# quick GPU check: selected tests + A/B timings. bash tools/gpu_quick.sh TAG "pytest args" [ab envs...]
TAG=$1; T=$2; shift 2
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
if [ -n "$T" ]; then timeout 1200 python -m pytest -x -q -p no:cacheprovider $T > gpurun_out/pytest_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_$TAG.log; fi
if [ $# -gt 0 ]; then bash tools/ab.sh $TAG "$@"; fi
echo done
