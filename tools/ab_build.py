"""Build an A/B variant of libczc.so with extra nvcc flags (development aid).

    python tools/ab_build.py NAME [-DFOO=1 ...]   ->  abtest/NAME.so
"""
import os, subprocess, sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
name, flags = sys.argv[1], sys.argv[2:]
os.makedirs(os.path.join(ROOT, "abtest"), exist_ok=True)
env = dict(os.environ, CZC_NVCC_EXTRA=" ".join(flags),
           CZC_OBJ_DIR=os.path.join(ROOT, "abtest", "obj_" + name),
           CZC_SO_OUT=os.path.join(ROOT, "abtest", name + ".so"))
subprocess.run([sys.executable, "-m", "paper_conf_cluster_yudgtc21_b200.build"], cwd=ROOT, env=env, check=True,
               stdout=subprocess.DEVNULL)
print(os.path.join("abtest", name + ".so"))
