#!/bin/bash
# Build libipt.so (forwarding to _build.py) and print errors / register use of matching kernels.
# usage: tools/build.sh [kernel-regex]
cd "$(dirname "$0")/.."
python -c "
import importlib.util
spec=importlib.util.spec_from_file_location('b','paper_conf_ppopp_catanzarokg14_b200/_build.py'); b=importlib.util.module_from_spec(spec); spec.loader.exec_module(b); b.build(verbose=True)" > /tmp/ipt_build.log 2>&1
rc=$?
grep -i "error" /tmp/ipt_build.log | sort | uniq | head -20
if [ -n "$1" ]; then grep -A2 "Compiling entry.*$1" /tmp/ipt_build.log | grep -E "Used|spill" | sort | uniq -c | head -20; fi
exit $rc
