"""Build an experiment copy of libac.so with extra nvcc defines (development
tool): python scripts/build_variant.py OUT.so -DAC_COOP_BATCH=2 ...
Objects go to build/obj_<name>; the in-tree libac.so is untouched."""
from __future__ import annotations

import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

from paper_conf_ipps_tranlhc13_b200 import _build  # noqa: E402


def main():
    out = Path(sys.argv[1]).resolve()
    defs = sys.argv[2:]
    obj_dir = ROOT / "build" / f"obj_{out.stem}"
    obj_dir.mkdir(parents=True, exist_ok=True)

    def one(src: Path) -> Path:
        obj = obj_dir / (src.name + ".o")
        subprocess.check_call([_build.nvcc(), *_build.CFLAGS, *defs, f"-I{_build.INCLUDE}", f"-I{_build.CSRC}", "-c",
                               str(src), "-o", str(obj)])
        return obj

    with ThreadPoolExecutor(8) as ex:
        objs = list(ex.map(one, _build.sources()))
    out.parent.mkdir(parents=True, exist_ok=True)
    subprocess.check_call([_build.nvcc(), *_build.ARCH, "-shared", "-o", str(out), *map(str, objs), "-ldl"])
    print(out)


if __name__ == "__main__":
    main()
