"""Build alternative libsgr.so variants (macro settings) into tools/alt/ in parallel."""
import sys
import os
from concurrent.futures import ThreadPoolExecutor
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_licqfsty16_b200 import _build  # noqa: E402

ALT = os.path.join(os.path.dirname(os.path.abspath(__file__)), "alt")


def one(spec):
    name, flags = spec.split("=", 1) if "=" in spec else (spec, "")
    extra = [f"-D{f}" for f in flags.split(",") if f]
    os.makedirs(ALT, exist_ok=True)
    _build.build_cuda(force=True, out=os.path.join(ALT, name + ".so"), extra=extra, tag="obj_" + name)
    return name


if __name__ == "__main__":
    # e.g.  w512b4=SGR_WIN=512,SGR_MINB=4
    with ThreadPoolExecutor(4) as ex:
        for n in ex.map(one, sys.argv[1:]):
            print("built", n)
