#!/bin/bash
# Build A/B variants of libganns.so into ab/ (each: full build with extra -D flags),
# then rebuild the default library.  Usage: tools/build_variants.sh name "-DFOO=0" [name "-D..."]...
set -e
cd "$(dirname "$0")/.."
mkdir -p ab
B='import importlib.util as u; s=u.spec_from_file_location("b","paper_conf_icde_yuwzqzl22_b200/_build.py"); b=u.module_from_spec(s); s.loader.exec_module(b); b.build(force=True)'
while [ $# -ge 2 ]; do
  GANNS_NVCC_EXTRA="$2" python -c "$B"
  cp paper_conf_icde_yuwzqzl22_b200/libganns.so "ab/libganns_$1.so"
  echo "built ab/libganns_$1.so ($2)"
  shift 2
done
python -c "$B"
echo "rebuilt default"
