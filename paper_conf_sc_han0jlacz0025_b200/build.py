"""Build libmako.so in-tree with nvcc for sm_100a (parallel per translation unit).

    python -m paper_conf_sc_han0jlacz0025_b200.build [-j N] [--force]
"""
import argparse
import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OBJ = os.path.join(HERE, "build_obj")
LIB = os.path.join(HERE, "libmako.so")
ROOT = os.path.dirname(HERE)

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-O2", "--expt-relaxed-constexpr",
         "-I" + os.path.join(ROOT, "include"), "-I" + CSRC]


def sources():
    return sorted(f for f in os.listdir(CSRC) if f.endswith(".cu") or f.endswith(".cpp"))


def headers_mtime():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith(".h") or f.endswith(".cuh")]
    hs.append(os.path.join(ROOT, "include", "mako.h"))
    return max(os.path.getmtime(h) for h in hs)


def _compile(src, force, verbose, obj_dir=None, defines=()):
    obj = os.path.join(obj_dir or OBJ, src + ".o")
    sp = os.path.join(CSRC, src)
    if not force and os.path.exists(obj) and os.path.getmtime(obj) > max(os.path.getmtime(sp), headers_mtime()):
        return obj, ""
    pre = []
    if defines:  # nvcc splits -D values at commas: variant defines go through a pre-included header
        hdr = os.path.join(obj_dir, "mako_variant.h")
        pre = ["--pre-include", hdr]
    cmd = [NVCC] + ARCH + FLAGS + pre + ["-c", sp, "-o", obj]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr}")
    return obj, r.stderr


def build(force=False, jobs=None, verbose=False, variant=None, defines=()):
    """variant: experiment build with extra -D defines into libmako_<variant>.so (selected by MAKO_LIB)."""
    obj_dir = OBJ if not variant else OBJ + "_" + variant
    lib = LIB if not variant else os.path.join(HERE, "libmako_%s.so" % variant)
    os.makedirs(obj_dir, exist_ok=True)
    if defines:
        txt = "".join("#define %s %s\n" % tuple((d.split("=", 1) + [""])[:2]) for d in defines)
        hdr = os.path.join(obj_dir, "mako_variant.h")
        if not os.path.exists(hdr) or open(hdr).read() != txt:
            open(hdr, "w").write(txt)
            force = True
    srcs = sources()
    jobs = jobs or max(1, os.cpu_count() or 1)
    objs, logs = [], {}
    with cf.ThreadPoolExecutor(jobs) as ex:
        futs = {ex.submit(_compile, s, force, verbose, obj_dir, defines): s for s in srcs}
        for f in cf.as_completed(futs):
            o, log = f.result()
            objs.append(o)
            logs[futs[f]] = log
    objs.sort()
    if force or not os.path.exists(lib) or os.path.getmtime(lib) < max(os.path.getmtime(o) for o in objs):
        cmd = [NVCC] + ARCH + ["-shared", "-o", lib] + objs + ["-lcudart"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("link failed:\n" + r.stderr)
    return lib, logs


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("-j", type=int, default=None)
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-v", action="store_true", help="ptxas -v register/smem report")
    ap.add_argument("--variant", default=None, help="experiment build name (libmako_<variant>.so)")
    ap.add_argument("-D", action="append", default=[], help="extra define for a variant build")
    a = ap.parse_args()
    lib, logs = build(a.force, a.j, a.v, a.variant, a.D)
    if a.v:
        for k in sorted(logs):
            sys.stdout.write(f"== {k}\n{logs[k]}")
    print(lib)
