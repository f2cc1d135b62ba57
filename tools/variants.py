"""Build experiment variants of libsepo.so (compile-time switches) into exp/ and time them.

  python tools/variants.py build NAME:-DFLAG=1,-DX=2 ...     (here, CPU: nvcc cross-compile)
  python tools/variants.py run CFG:RATIO[:SCALE] ... -- NAME ...  (GPU box: time_job per variant)
The default library is the variant named 'base'. Results go to stdout as JSON lines.
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def build(specs):
    from tools.build import build_sepo
    os.makedirs(os.path.join(ROOT, "exp"), exist_ok=True)
    for spec in specs:
        name, _, flags = spec.partition(":")
        extra = [f for f in flags.split(",") if f]
        build_sepo(force=True, target=os.path.join(ROOT, "exp", f"lib_{name}.so"), extra=extra)


def run(jobs, names):
    for name in names:
        # NAME or NAME+VAR=VALUE[+VAR=VALUE]: library exp/lib_NAME.so with extra environment
        base, *envs = name.split("+")
        lib = os.path.join(ROOT, "exp", f"lib_{base}.so")
        env = dict(os.environ, SEPO_LIB=lib)
        env.update(dict(e.split("=", 1) for e in envs))
        for j in jobs:
            parts = j.split(":")
            cmd = [sys.executable, os.path.join(ROOT, "tools", "time_job.py")] + parts
            r = subprocess.run(cmd, env=env, capture_output=True, text=True, cwd=ROOT, timeout=600)
            line = (r.stdout.strip().splitlines() or ["{}"])[-1]
            try:
                d = json.loads(line)
            except Exception:
                d = {"error": (r.stderr or r.stdout)[-400:]}
            d["variant"] = name
            print(json.dumps(d), flush=True)


if __name__ == "__main__":
    if sys.argv[1] == "build":
        build(sys.argv[2:])
    else:
        i = sys.argv.index("--")
        run(sys.argv[2:i], sys.argv[i + 1:])
