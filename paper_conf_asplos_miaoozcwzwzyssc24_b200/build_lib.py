"""Builds libspecinfer.so in-tree with nvcc for sm_100a (B200) only.

    python -m paper_conf_asplos_miaoozcwzwzyssc24_b200.build_lib [--force] [--verbose]
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
import tempfile

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libspecinfer.so")
DEBUG_LIB = os.path.join(HERE, "libspecinfer_debug.so")   # -DSPECINFER_DEBUG_HOOKS (tools only)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2", "--expt-relaxed-constexpr",
         "-I", os.path.join(ROOT, "include")]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale(lib=LIB) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "specinfer.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, extra=(), debug_hooks: bool = False, out=None) -> str:
    """Compiles every csrc/*.cu for sm_100a and links libspecinfer.so; with debug_hooks, the
    development variant libspecinfer_debug.so (pipeline traces, experiment switches); with `out`,
    an A/B variant at that path (development tools: `extra` holds its -D switches)."""
    target = out or (DEBUG_LIB if debug_hooks else LIB)
    if debug_hooks:
        extra = tuple(extra) + ("-DSPECINFER_DEBUG_HOOKS",)
    if not force and not _stale(target):
        return target
    with tempfile.TemporaryDirectory() as td:
        objs = []
        procs = []
        for src in sources():
            obj = os.path.join(td, os.path.basename(src) + ".o")
            cmd = [NVCC, *ARCH, *FLAGS, *extra, "-c", src, "-o", obj]
            if verbose:
                cmd.insert(1, "-Xptxas=-v")
                print(" ".join(cmd), flush=True)
            procs.append((src, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
            objs.append(obj)
        failed = False
        for src, pr in procs:
            out, _ = pr.communicate()
            if pr.returncode != 0 or verbose:
                sys.stderr.write(out.decode(errors="replace"))
            if pr.returncode != 0:
                failed = True
                sys.stderr.write(f"nvcc failed on {src}\n")
        if failed:
            raise RuntimeError("libspecinfer build failed")
        tmp = target + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart_static", "-lrt", "-ldl",
                               "-lpthread"])
        os.replace(tmp, target)
    return target


if __name__ == "__main__":
    # python -m ...build_lib [--force] [--verbose] [--debug-hooks] [--out PATH -DNAME ...]
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
    print(build(force="--force" in sys.argv or out is not None, verbose="--verbose" in sys.argv,
                debug_hooks="--debug-hooks" in sys.argv, out=out,
                extra=tuple(a for a in sys.argv[1:] if a.startswith("-D"))))
