#!/bin/bash
for r in 1 2 3; do for pk in "$@"; do echo -n "$pk "; GALLATIN_PKG_ROOT=$PWD/$pk timeout 300 python tools/mixed_probe.py 2>/dev/null | head -2 | tr '\n' ' '; echo; done; done
