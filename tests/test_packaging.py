"""Packaging checks that need no GPU."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_libmm_then_torch_import():
    # libmm.so must not pin a second NCCL build: torch has to import after it.
    code = "import paper_conf_icpp_shenvms15_b200.mm as m; import torch, torch.distributed; print('ok')"
    p = subprocess.run([sys.executable, "-c", code], cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert p.returncode == 0 and "ok" in p.stdout, p.stderr


def test_no_link_time_cuda_driver_or_nccl():
    out = subprocess.run(["ldd", os.path.join(ROOT, "paper_conf_icpp_shenvms15_b200", "libmm.so")],
                         capture_output=True, text=True).stdout
    assert "libnccl" not in out and "libcuda.so" not in out


def test_product_package_does_not_import_oracle():
    # the product path must never route through the oracle
    pkg = os.path.join(ROOT, "paper_conf_icpp_shenvms15_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                # comments may cite the oracle; code may not name its module or library
                code = "\n".join(ln.split("//")[0].split("#")[0] for ln in src.split("\n"))
                assert "oracle" not in code, f
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "or_stream" not in src and "_numeric" not in src, f
