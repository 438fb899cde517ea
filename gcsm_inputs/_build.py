"""Build libgcsm_inputs.so (plain g++ + OpenMP; no GPU code)."""
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libgcsm_inputs.so")


def build(force: bool = False) -> str:
    src = os.path.join(HERE, "gen.cpp")
    if not force and os.path.exists(LIB_PATH) and os.path.getmtime(LIB_PATH) >= os.path.getmtime(src):
        return LIB_PATH
    cmd = ["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-fopenmp", src, "-o", LIB_PATH + ".tmp"]
    subprocess.check_call(cmd)
    os.replace(LIB_PATH + ".tmp", LIB_PATH)
    return LIB_PATH
