"""Build compile-time tuning variants of libgpumem.so into exp/<name>/ (travels to the GPU box).
    python tools/variants.py name=-DA=1,-DB=2 [name2=...]
Then run any tool with GPUMEM_LIB=exp/<name>/libgpumem.so."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_abu_dolehkac14_b200 import _build
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
for arg in sys.argv[1:]:
    name, _, defs = arg.partition('=')
    d = os.path.join(root, 'exp', name)
    os.makedirs(d, exist_ok=True)
    lib = _build.build(lib=os.path.join(d, 'libgpumem.so'), objdir=os.path.join(root, 'build', 'variants', name),
                       defines=[x for x in defs.split(',') if x])
    print(lib, flush=True)
