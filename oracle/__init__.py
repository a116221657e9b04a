"""CPU ORACLE for the ParSecureML hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything under ``oracle/``.  The product package
``paper_conf_icpp_chenzzzz020_b200`` never imports it, and this package never imports the
product package: the two share no code.  The only module both sides use is ``synth`` (seeded
plaintext input generators, none of the method's arithmetic).

Layout:
  psml_oracle.c  plain C simulation of both parties in uint64 wraparound (PRG, encode, share,
                 dealer, Beaver matmul/Hadamard, truncation, secure MSB, CSR delta codec)
  core.py        ctypes marshalling of psml_oracle.c + im2col + ReLU/Eq. 9 assembly
  protocol.py    the training / inference protocols of PAPER.md Sec. 4.3 (L199-L207) for
                 linear/logistic regression, MLP and CNN, with the call-id layout of DESIGN.md
  plain.py       plaintext fp64 numpy training (the 2^-12 weight pin of BASELINE north_star)
  bruteforce.py  pure-Python big-integer definitions for tiny inputs (pins for the C oracle)

Parity status per function is listed in DESIGN.md ("Oracle pins").  Functions without an
independent pin say "parity unpinned" in their docstring.
"""
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
SRC_PATH = os.path.join(_HERE, "psml_oracle.c")


def build(force: bool = False) -> str:
    """Compile psml_oracle.c with gcc -O2 -fopenmp into oracle/liboracle.so."""
    if (not force and os.path.exists(LIB_PATH)
            and os.path.getmtime(LIB_PATH) >= os.path.getmtime(SRC_PATH)):
        return LIB_PATH
    cmd = ["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11", "-Wall",
           "-fvisibility=hidden", "-o", LIB_PATH + ".tmp", SRC_PATH, "-lm"]
    subprocess.check_call(cmd)
    os.replace(LIB_PATH + ".tmp", LIB_PATH)
    return LIB_PATH
