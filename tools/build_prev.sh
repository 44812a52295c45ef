#!/bin/bash
# build the committed HEAD (or $1) as variant "prev" for tools/ab.sh
REV=${1:-HEAD}
rm -rf /tmp/prev_src && mkdir -p /tmp/prev_src && git archive $REV paper_conf_isca_stephensonhlejn15_b200/csrc | tar -x -C /tmp/prev_src
python tools/build_variant.py prev --src=/tmp/prev_src/paper_conf_isca_stephensonhlejn15_b200/csrc 2>&1 | grep -v "warning"
