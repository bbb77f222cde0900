#!/bin/bash
# build + CPU test suite; run before every GPU call
cd "$(dirname "$0")/.." && python -c "import __graft_entry__ as g; g.build_cuda(); g.build_cpu()" && timeout 900 python -m pytest tests -q -m "not gpu" -x 2>&1 | tail -1
