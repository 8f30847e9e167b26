"""Compile the plain-C oracle ``oracle/liblfd_ref.so`` (test infrastructure only).

Flags: -O2 -ffp-contract=off (no FMA contraction, so the oracle's roundoff is that of the literal
formulas) and -fcx-limited-range (textbook complex multiply, no Annex-G NaN recovery calls).
"""
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "lfd_ref.c")
LIB = os.path.join(HERE, "liblfd_ref.so")


def build(force: bool = False) -> str:
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= os.path.getmtime(SRC):
        return LIB
    cmd = ["gcc", "-std=c11", "-O2", "-ffp-contract=off", "-fcx-limited-range", "-fPIC", "-shared",
           "-Wall", "-Wextra", "-o", LIB + ".tmp", SRC, "-lm"]
    subprocess.run(cmd, check=True)
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    print(build(force=True))
