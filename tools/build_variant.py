"""Build an A/B variant of libmobius.so with extra nvcc defines for one
source file (kernel tuning knobs), e.g.
  python tools/build_variant.py flash.cu MOBIUS_FLASH_POLY_PAIRS=0 -> tools/gpu/var/libmobius_<tag>.so
then time it with MOBIUS_LIB_PATH=<that .so> python tools/flash_time.py."""
import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import importlib.util  # noqa: E402

spec = importlib.util.spec_from_file_location("b", os.path.join(ROOT, "paper_conf_asplos_fengxtwls23_b200", "build.py"))
b = importlib.util.module_from_spec(spec)
spec.loader.exec_module(b)


def main():
    src, defs = sys.argv[1], sys.argv[2:]
    tag = "_".join(d.replace("=", "") for d in defs) or "base"
    out_dir = os.path.join(ROOT, "tools", "gpu", "var")
    os.makedirs(out_dir, exist_ok=True)
    b.build()
    objs = sorted(glob.glob(os.path.join(b.BUILD, "*.o")))
    vobj = os.path.join(out_dir, f"{src}.{tag}.o")
    cmd = [b.NVCC] + b.ARCH + b.NVFLAGS + [f"-D{d}" for d in defs] + ["-c", os.path.join(b.CSRC, src), "-o", vobj]
    subprocess.check_call(cmd)
    objs = [o for o in objs if os.path.basename(o) != src + ".o"] + [vobj]
    lib = os.path.join(out_dir, f"libmobius_{tag}.so")
    subprocess.check_call([b.NVCC] + b.ARCH + ["-shared", "-o", lib] + objs + ["-lcudart", "-ldl", "-lpthread"])
    print(lib)


if __name__ == "__main__":
    main()
