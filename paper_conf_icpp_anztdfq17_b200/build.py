"""Build libbj.so (the CUDA path, sm_100a) in-tree with nvcc.

Every kernel translation unit is compiled for ``sm_100a`` only
(``-gencode arch=compute_100a,code=sm_100a``) with ``-lineinfo`` and IEEE
arithmetic flags (no fast math: ``-ftz=false -prec-div=true``).  The GETRF /
GETRS kernels are instantiated per (dtype, size class) in separate objects so
they compile in parallel.  ``python -m paper_conf_icpp_anztdfq17_b200.build``.
"""
from __future__ import annotations

import concurrent.futures as cf
import hashlib
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(ROOT, "include")
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libbj.so")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-ftz=false", "-prec-div=true",
         "-prec-sqrt=true", "-fmad=true", "-Xptxas", "-v", "-I", INCLUDE, "-I", CSRC]

CLASSES = [(1, 4), (5, 8), (9, 16), (17, 32)]
DTYPES = ["double", "float"]


def _jobs():
    jobs = []
    for src in ("api.cu", "layout.cu", "getrf.cu", "getrs.cu", "extract.cu", "synth.cu", "supervar.cu", "getri.cu", "selftest.cu", "krylov.cu"):
        jobs.append((src, [], src.replace(".cu", ".o")))
    for kind in ("getrf", "getrs"):
        for dt in DTYPES:
            classes = CLASSES if kind == "getrs" else CLASSES[:3] + [(m, m) for m in range(17, 33)]
            for lo, hi in classes:
                jobs.append((f"{kind}_inst.cu", [f"-DBJ_R={dt}", f"-DBJ_LO={lo}", f"-DBJ_HI={hi}"],
                             f"{kind}_{dt[0]}_{lo}_{hi}.o"))
    return jobs


def _sources_digest():
    h = hashlib.sha256()
    for d in (CSRC, INCLUDE):
        for f in sorted(os.listdir(d)):
            if f.endswith((".cu", ".cuh", ".h")):
                h.update(f.encode())
                with open(os.path.join(d, f), "rb") as fh:
                    h.update(fh.read())
    h.update(" ".join(ARCH + FLAGS).encode())
    return h.hexdigest()


def _headers_digest():
    h = hashlib.sha256()
    for d in (CSRC, INCLUDE):
        for f in sorted(os.listdir(d)):
            if f.endswith((".cuh", ".h")):
                h.update(f.encode())
                with open(os.path.join(d, f), "rb") as fh:
                    h.update(fh.read())
    return h.hexdigest()


def _job_digest(job, headers):
    src, defs, _ = job
    h = hashlib.sha256()
    h.update(headers.encode())
    h.update(" ".join(ARCH + FLAGS + defs).encode())
    with open(os.path.join(CSRC, src), "rb") as fh:
        h.update(fh.read())
    return h.hexdigest()


def _compile(job, headers=None):
    """Compile one object unless its sources (file + every header + flags)
    are unchanged since the last build of that object."""
    src, defs, obj = job
    out = os.path.join(BUILD, obj)
    stamp = out + ".digest"
    dg = _job_digest(job, headers or _headers_digest())
    if os.path.exists(out) and os.path.exists(stamp) and open(stamp).read() == dg:
        log = out + ".log"
        return obj, open(log).read() if os.path.exists(log) else ""
    cmd = [NVCC, *ARCH, *FLAGS, *defs, "-c", os.path.join(CSRC, src), "-o", out]
    p = subprocess.run(cmd, capture_output=True, text=True)
    if p.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src} {defs}:\n{p.stderr[-4000:]}")
    with open(out + ".log", "w") as fh:
        fh.write(p.stderr)
    with open(stamp, "w") as fh:
        fh.write(dg)
    return obj, p.stderr


def build(force: bool = False, jobs: int | None = None, verbose: bool = False) -> str:
    """Compile (if sources changed) and link libbj.so; returns its path."""
    os.makedirs(BUILD, exist_ok=True)
    digest = _sources_digest()
    stamp = os.path.join(BUILD, "digest")
    if not force and os.path.exists(LIB) and os.path.exists(stamp) and open(stamp).read() == digest:
        return LIB
    todo = _jobs()
    n = jobs or min(len(todo), os.cpu_count() or 4)
    logs = []
    headers = _headers_digest()
    with cf.ThreadPoolExecutor(max_workers=n) as ex:
        for obj, log in ex.map(lambda j: _compile(j, headers), todo):
            logs.append(f"== {obj}\n{log}")
    with open(os.path.join(BUILD, "ptxas.log"), "w") as fh:
        fh.write("\n".join(logs))
    objs = [os.path.join(BUILD, o) for _, _, o in todo]
    tmp = LIB + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart_static", "-lrt", "-ldl", "-lpthread"]
    p = subprocess.run(cmd, capture_output=True, text=True)
    if p.returncode != 0:
        raise RuntimeError(f"link failed:\n{p.stderr[-4000:]}")
    os.replace(tmp, LIB)
    with open(stamp, "w") as fh:
        fh.write(digest)
    if verbose:
        print("\n".join(logs))
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
