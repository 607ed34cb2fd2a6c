"""Loaders for the hand-counted fixtures in tests/golden/ (each file cites its source)."""
import ast
import os

HERE = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_corpus(name):
    docs, terms, hdr = [], {}, {}
    for line in open(os.path.join(HERE, name), encoding="utf-8"):
        line = line.rstrip("\n")
        if not line or line.startswith("#"):
            continue
        key, rest = line.split(" ", 1)
        if key == "doc":
            docs.append(ast.literal_eval(rest))
        elif key == "term":
            lit_end = rest.index('"', 2) + 1
            term = ast.literal_eval(rest[:lit_end])
            fields = rest[lit_end:].split()
            df, cf = int(fields[0]), int(fields[1])
            posts = [tuple(int(x) for x in p.split(":")) for p in fields[2:]]
            assert len(posts) == df and sum(t for _, t in posts) == cf, name
            terms[term] = posts
        else:
            hdr[key] = int(rest)
    return docs, hdr, terms


def load_buckets():
    out = []
    for line in open(os.path.join(HERE, "table1_buckets.txt"), encoding="utf-8"):
        if line.startswith("b"):
            parts = line.split()
            out.append((ast.literal_eval(parts[0]), int(parts[1]), " ".join(parts[2:])))
    return out
