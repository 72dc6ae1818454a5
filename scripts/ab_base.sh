#!/bin/bash
# Build the committed HEAD library into ab/librgsqr_base.so (A/B baseline; RGSQR_LIB=ab/librgsqr_base.so selects it).
set -e
cd "$(dirname "$0")/.."
rm -rf /tmp/ab_src && mkdir -p /tmp/ab_src ab
git archive HEAD paper_conf_icpp_zhangw21_b200 include | tar -x -C /tmp/ab_src
python -c "import sys; sys.path.insert(0, '/tmp/ab_src'); from paper_conf_icpp_zhangw21_b200 import build; print(build.build(force=True))"
cp /tmp/ab_src/paper_conf_icpp_zhangw21_b200/librgsqr.so ab/librgsqr_base.so
