#!/bin/bash
# Build libsgr.so with extra nvcc flags into tools/alt/<name>.so, then rebuild the default.
set -e
cd "$(dirname "$0")/.."
name=$1; shift
NVCC_APPEND_FLAGS="$*" python -c "from paper_conf_ipps_licqfsty16_b200 import _build; _build.build_cuda(force=True)" > /tmp/build_$name.log 2>&1 || { tail -20 /tmp/build_$name.log; exit 1; }
mkdir -p tools/alt && cp paper_conf_ipps_licqfsty16_b200/lib/libsgr.so tools/alt/$name.so
python -c "from paper_conf_ipps_licqfsty16_b200 import _build; _build.build_cuda(force=True)" > /tmp/build_default.log 2>&1 || { tail -20 /tmp/build_default.log; exit 1; }
echo "built tools/alt/$name.so and the default lib"
