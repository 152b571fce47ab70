"""Build a variant of libmcl.so for A/B timing (scripts/ab_lib.py): the listed sources
recompiled with extra nvcc flags (e.g. -DMCL_BATCH_MINB=3), linked with the in-tree objects.

    python scripts/build_variant.py ab/libmcl_v1.so search_batch.cu -DMCL_BATCH_MINB=3
"""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_ajipbf15_b200 import build as B  # noqa: E402


def main():
    out, src, flags = sys.argv[1], sys.argv[2].split(","), sys.argv[3:]
    B.build()
    os.makedirs(os.path.dirname(os.path.abspath(out)), exist_ok=True)
    tag = os.path.splitext(os.path.basename(out))[0]
    objs = []
    for s in B.SOURCES:
        obj = os.path.join(B.BUILD, s + ".o")
        if s in src:
            obj = os.path.join(B.BUILD, f"{s}.{tag}.o")
            cmd = [B.NVCC] + B._flags() + flags + ["-c", os.path.join(B.CSRC, s), "-o", obj]
            r = subprocess.run(cmd, capture_output=True, text=True)
            if r.returncode:
                sys.exit(" ".join(cmd) + "\n" + r.stderr)
        objs.append(obj)
    r = subprocess.run([B.NVCC] + B.ARCH + ["-shared", "-o", out] + objs + ["-ldl", "-lpthread"],
                       capture_output=True, text=True)
    if r.returncode:
        sys.exit(r.stderr)
    print(out)


if __name__ == "__main__":
    main()
