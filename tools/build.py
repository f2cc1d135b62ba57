"""In-tree build of every native library (sm_100a CUDA + host C++).

  paper_conf_ipps_mokhtaris17_b200/lib/libsepo.so   — the product: C-ABI SEPO hash table (CUDA)
  gen/libsepogen.so                                  — synthetic input generators (host + device)
  oracle/liboracle.so                                — CPU oracle (test infrastructure; plain C++)

Run `python tools/build.py` (or `__graft_entry__.build()`). Rebuilds only what is stale.
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
PKG = os.path.join(ROOT, "paper_conf_ipps_mokhtaris17_b200")


def _nccl_dirs():
    try:
        import nvidia.nccl  # noqa: F401
        base = list(nvidia.nccl.__path__)[0]
        return os.path.join(base, "include"), os.path.join(base, "lib")
    except Exception:
        return None, None


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def _run(cmd):
    print("+", " ".join(cmd), flush=True)
    subprocess.check_call(cmd, cwd=ROOT)


def _files(d, exts):
    out = []
    for dp, _, fns in os.walk(d):
        for f in fns:
            if os.path.splitext(f)[1] in exts:
                out.append(os.path.join(dp, f))
    return sorted(out)


def build_gen(force=False):
    tgt = os.path.join(ROOT, "gen", "libsepogen.so")
    deps = _files(os.path.join(ROOT, "gen"), {".h", ".cpp", ".cu"})
    if not force and not _stale(tgt, deps):
        return tgt
    _run([NVCC, "-O3", "-std=c++17", *ARCH, "-shared", "-Xcompiler", "-fPIC,-fopenmp", "-lineinfo",
          "gen/gen_dev.cu", "gen/gen_host.cpp", "-lgomp", "-o", tgt])
    return tgt


def build_oracle(force=False):
    tgt = os.path.join(ROOT, "oracle", "liboracle.so")
    deps = _files(os.path.join(ROOT, "oracle"), {".h", ".cpp"})
    if not force and not _stale(tgt, deps):
        return tgt
    _run(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "oracle/oracle.cpp", "-o", tgt])
    return tgt


def build_sepo(force=False, target=None, extra=()):
    os.makedirs(os.path.join(PKG, "lib"), exist_ok=True)
    tgt = target or os.path.join(PKG, "lib", "libsepo.so")
    csrc = os.path.join(PKG, "csrc")
    deps = _files(csrc, {".h", ".cuh", ".cu", ".cpp"}) + _files(os.path.join(ROOT, "include"), {".h"})
    if not force and not _stale(tgt, deps):
        return tgt
    srcs = [os.path.relpath(f, ROOT) for f in _files(csrc, {".cu", ".cpp"})]
    inc, lib = _nccl_dirs()
    cmd = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", "-shared", "-Xcompiler", "-fPIC,-pthread",
           "-Xptxas", "-v" if os.environ.get("SEPO_PTXAS_V") else "-O3",
           "-Iinclude", "-I" + os.path.relpath(csrc, ROOT)]
    if inc:
        cmd += ["-I" + inc, "-DSEPO_WITH_NCCL=1", "-L" + lib, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + lib]
    cmd += list(extra) + srcs + ["-o", tgt]
    _run(cmd)
    return tgt


def build_all(force=False):
    return [build_gen(force), build_oracle(force), build_sepo(force)]


if __name__ == "__main__":
    force = "--force" in sys.argv
    which = [a for a in sys.argv[1:] if not a.startswith("--")]
    fns = {"gen": build_gen, "oracle": build_oracle, "sepo": build_sepo}
    if not which:
        build_all(force)
    else:
        for w in which:
            fns[w](force)
