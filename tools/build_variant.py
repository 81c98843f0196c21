"""Build an experiment variant of libflep.so with extra nvcc flags into build_variants/<name>.so
(flep.py loads it with FLEP_LIB_PATH=...). Usage: python tools/build_variant.py name -DX=1 ..."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_wulzj17_b200 import build as B  # noqa: E402


def main():
    name, extra = sys.argv[1], sys.argv[2:]
    os.makedirs(os.path.join(ROOT, "build_variants"), exist_ok=True)
    out = os.path.join(ROOT, "build_variants", name + ".so")
    cmd = [B._nvcc()] + B.NVCC_FLAGS + extra + ["-o", out] + B.sources() + ["-lpthread"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode:
        sys.exit(r.stdout + r.stderr)
    print(out)


if __name__ == "__main__":
    main()
