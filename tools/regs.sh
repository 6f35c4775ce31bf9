#!/bin/bash
# registers / stack per J/K kernel of an in-tree build: tools/regs.sh [libmako.so] [pattern]
lib=${1:-paper_conf_sc_han0jlacz0025_b200/libmako.so}
cuobjdump -res-usage "$lib" 2>/dev/null | awk '/Function/{f=$2} /REG:/{match($0,/REG:[0-9]+/); r=substr($0,RSTART,RLENGTH); match($0,/STACK:[0-9]+/); s=substr($0,RSTART,RLENGTH); match($0,/SHARED:[0-9]+/); sh=substr($0,RSTART,RLENGTH); print f, r, s, sh}' | sed 's/_ZN4mako//; s/EENS_6JKArgsE:*//; s/ILi/</; s/ELi/,/; s/E</</' | grep -E "${2:-jk|slab|kf|tpq}"
