"""The boundary used from plain C: examples/c_abi_parity.c links libfeves_me.so and the
C oracle, runs INT / ME / SME through include/feves_me.h and checks bit-exactness."""
import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_c_program_through_the_c_abi(tmp_path):
    import __graft_entry__ as g
    g.build()
    exe = str(tmp_path / "c_abi_parity")
    cuda = "/usr/local/cuda"
    subprocess.check_call(["gcc", "-O2", "-I", os.path.join(ROOT, "include"), "-I", f"{cuda}/include", "-o", exe,
                           os.path.join(ROOT, "examples", "c_abi_parity.c"),
                           "-L", os.path.join(ROOT, "paper_conf_icpp_ilicmrs14_b200"), "-lfeves_me",
                           "-L", os.path.join(ROOT, "oracle"), "-loracle", "-L", f"{cuda}/lib64", "-lcudart"])
    env = dict(os.environ)
    env["LD_LIBRARY_PATH"] = ":".join([os.path.join(ROOT, "paper_conf_icpp_ilicmrs14_b200"),
                                       os.path.join(ROOT, "oracle"), f"{cuda}/lib64",
                                       env.get("LD_LIBRARY_PATH", "")])
    out = subprocess.run([exe], capture_output=True, text=True, env=env, timeout=300)
    assert out.returncode == 0, out.stdout + out.stderr
    assert "bit-exact" in out.stdout
