"""Force-rebuild libsq.so with extra nvcc defines (experiments): python tools/build_variant.py -DFOO=1 ..."""
import importlib.util
import os
import sys

os.environ["SQ_NVCC_EXTRA"] = " ".join(sys.argv[1:])
spec = importlib.util.spec_from_file_location(
    "b", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_cluster_zhaowplw25_b200", "build.py"))
m = importlib.util.module_from_spec(spec)
spec.loader.exec_module(m)
m.build(force=True)
print("built with", os.environ["SQ_NVCC_EXTRA"])
