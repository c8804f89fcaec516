"""Build the C-ABI library ``libplr_b200.so`` in-tree with nvcc for sm_100a.

Every .cu/.cpp under csrc/ is compiled in parallel with
``-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo`` (fp32 kernels with
``-ftz=true``: denormals flushed as in the paper) and linked into
one shared library with the static CUDA runtime.  No torch types cross the
library boundary; the Python binding loads it with ctypes.
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
# experiment variants: PLR_VARIANT="name:S.D.NL[.X.W]:S.D.NL[.X.W][:DEFS]" (DECAY config,
# generic config, extra defines joined by '+') builds libplr_b200_<name>.so
_VAR = os.environ.get("PLR_VARIANT")
_SUFFIX = "" if not _VAR else "_" + _VAR.split(":")[0]
BUILD = os.path.join(HERE, "_build" + _SUFFIX)
LIB = os.path.join(HERE, "libplr_b200%s.so" % _SUFFIX)
INCLUDE = os.path.join(os.path.dirname(HERE), "include")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-I" + INCLUDE, "-I" + CSRC,
          "--ftz=true", "--prec-div=true", "--prec-sqrt=true", "--fmad=true"]
if _VAR:   # name:S.D.NL:S.D.NL[:extra -D defines separated by +]  (nvcc splits -D values on ',')
    _p = _VAR.split(":")
    for _tag, _cfg in (("DEC", _p[1]), ("GEN", _p[2])):
        _v = _cfg.split(".") + ["15", "8", "3" if _tag == "DEC" else "2"][len(_cfg.split(".")) - 3:]
        for _name, _val in zip(("S", "D", "NL", "X", "W", "MINB"), _v):
            COMMON += ["-DPLR_%s_%s=%s" % (_tag, _name, _val)]
    if len(_p) > 3:
        COMMON += ["-D" + d for d in _p[3].split("+") if d]


def _sources():
    return sorted(f for f in os.listdir(CSRC) if f.endswith((".cu", ".cpp")))


def _headers_mtime():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    hs.append(os.path.join(INCLUDE, "plr.h"))
    return max(os.path.getmtime(h) for h in hs)


def _compile(src, verbose):
    obj = os.path.join(BUILD, src + ".o")
    path = os.path.join(CSRC, src)
    if os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(path), _headers_mtime()):
        return obj, ""
    cmd = [NVCC] + ARCH + COMMON + ["-c", path, "-o", obj]
    if src.endswith(".cpp"):
        cmd = [NVCC] + COMMON + ["-x", "c++", "-c", path, "-o", obj]
    if verbose and src.endswith(".cu"):
        cmd.insert(1, "-Xptxas=-v")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, " ".join(cmd), r.stderr))
    return obj, r.stderr


def build(verbose: bool = False, force: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    if force:
        for f in os.listdir(BUILD):
            os.remove(os.path.join(BUILD, f))
    srcs = _sources()
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        results = list(ex.map(lambda s: _compile(s, verbose), srcs))
    objs = [o for o, _ in results]
    if verbose:
        for (o, log), s in zip(results, srcs):
            if log:
                sys.stderr.write("== %s ==\n%s\n" % (s, log))
    newest = max(os.path.getmtime(o) for o in objs)
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < newest:
        tmp = LIB + ".tmp%d" % os.getpid()
        cmd = [NVCC] + ARCH + ["-shared", "-o", tmp] + objs + ["-ldl", "-cudart", "static"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n%s\n%s" % (" ".join(cmd), r.stderr))
        os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(verbose="-v" in sys.argv, force="-f" in sys.argv))
