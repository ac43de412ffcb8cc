#!/bin/bash
# Build libpsb.so of git revision $1 into paper_conf_icpp_namkn16_b200/libpsb_$2.so (A/B timing).
set -e
REV=$1; TAG=$2; WT=/tmp/psb_wt_$TAG
rm -rf $WT; git -C /root/repo worktree prune; git -C /root/repo worktree add -f $WT $REV >/dev/null
make -C $WT/paper_conf_icpp_namkn16_b200/csrc -j8 OUT=/root/repo/paper_conf_icpp_namkn16_b200/libpsb_$TAG.so OBJDIR=/tmp/psb_obj_$TAG >/dev/null 2>&1
git -C /root/repo worktree remove --force $WT
echo built /root/repo/paper_conf_icpp_namkn16_b200/libpsb_$TAG.so
