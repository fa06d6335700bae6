"""Diagnostic: time COLOR-Deg2 / COLOR-NONE for several libsym builds ($SYM_LIB) x JP modes."""
import os, subprocess, sys
HERE = os.path.dirname(os.path.abspath(__file__))
scale = sys.argv[1]
modes = os.environ.get("MODES", "levels").split(",")
kinds = os.environ.get("KINDS", "degk:2").split(",")
for lib in sys.argv[2:]:
    for kind in kinds:
        k, p = kind.split(":")
        for mode in modes:
            env = dict(os.environ, SYM_JP_MODE=mode, SYM_LIB=os.path.abspath(lib))
            print("lib", os.path.basename(lib), end=" ", flush=True)
            subprocess.run([sys.executable, os.path.join(HERE, "jp_modes.py"), "child", scale, k, p], env=env, timeout=900)
