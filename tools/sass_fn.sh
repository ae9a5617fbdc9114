#!/bin/bash
# dump the SASS of one kernel of libskipper.so: tools/sass_fn.sh NAME_SUBSTRING
cuobjdump -sass paper_conf_micro_singhslsknnd22_b200/libskipper.so | awk -v pat="$1" '
  /Function :/ { on = index($0, pat) > 0 }
  on { print }'
